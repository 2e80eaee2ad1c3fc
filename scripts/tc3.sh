# brute (persistent tcgen05) + projection check: parity tests, c5 bench
mkdir -p gpurun_out
T=${1:-tc3}
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
timeout 400 python -m pytest tests/test_gpu_brute_tc.py tests/test_gpu_project.py tests/test_gpu_parity.py -k "brute or project" -x -q > gpurun_out/${T}_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/${T}_pytest.txt
tail -15 gpurun_out/${T}_pytest.txt
timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/${T}_c5.json 2> gpurun_out/${T}_c5.err; echo "bench rc=$?"
tail -3 gpurun_out/${T}_c5.err
python -c "import json;d=json.loads([l for l in open('gpurun_out/${T}_c5.json') if l.startswith('{')][-1]);print(d['value'],d['kernels_us'],d['roofline'])"
