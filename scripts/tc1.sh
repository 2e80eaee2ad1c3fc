mkdir -p gpurun_out
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
timeout 300 python -m pytest tests/test_gpu_brute_tc.py tests/test_gpu_parity.py -k brute -x -q > gpurun_out/tc1_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/tc1_pytest.txt
tail -30 gpurun_out/tc1_pytest.txt
timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/tc1_c5.json 2> gpurun_out/tc1_c5.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/tc1_c5.json; tail -3 gpurun_out/tc1_c5.err
SS_BRUTE_POPC=1 timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/tc1_c5_popc.json 2>&1; echo "popc rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/tc1_c5_popc.json').read().strip().splitlines()[-1]);print(d['value'],d['kernels_us'])"
