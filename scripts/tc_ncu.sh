# full ncu capture of the brute kernels (c5 workload)
mkdir -p gpurun_out
T=${1:-tcn}
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"brute_tc_kernel" -s 2 -c 1 -o gpurun_out/${T}_prof -f python bench.py --config c5 --steps 3 --warmup 3 --ring 4 --no-cpu-baseline --inflight 1 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu full rc=$?"
tail -2 gpurun_out/${T}_ncu.log
