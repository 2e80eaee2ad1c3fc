# brute matcher check: parity tests, c5 bench, ncu launch list + full capture of the brute kernels
mkdir -p gpurun_out
T=${1:-tc2}
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
timeout 300 python -m pytest tests/test_gpu_brute_tc.py tests/test_gpu_parity.py -k brute -x -q > gpurun_out/${T}_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/${T}_pytest.txt
tail -3 gpurun_out/${T}_pytest.txt
timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/${T}_c5.json 2> gpurun_out/${T}_c5.err; echo "bench rc=$?"
python -c "import json;d=json.loads([l for l in open('gpurun_out/${T}_c5.json') if l.startswith('{')][-1]);print(d['value'],d['kernels_us'],d['roofline'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_c5.csv python bench.py --config c5 --steps 4 --warmup 3 --ring 8 --no-cpu-baseline --inflight 1 > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"brute" -s 6 -c 3 -o gpurun_out/${T}_prof_c5 -f python bench.py --config c5 --steps 4 --warmup 3 --ring 8 --no-cpu-baseline --inflight 1 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu full rc=$?"
tail -3 gpurun_out/${T}_ncu.log
