# c2 throughput vs ticks in flight
mkdir -p gpurun_out
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
for P in 1 2 4 6 8 12; do
  timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --inflight $P > gpurun_out/sweep_if$P.json 2>/dev/null
  python -c "import json;d=json.loads([l for l in open('gpurun_out/sweep_if$P.json') if l.startswith('{')][-1]);print($P, round(d['value']), d['latency_ms']['p50'], round(d['e2e']['value']))"
done
