set -u
OUT=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for C in c1 c4; do
  timeout 600 python bench.py --config $C --steps 100 --warmup 5 --no-cpu-baseline > $OUT/bench_r02h_$C.json 2> $OUT/bench_r02h_$C.err
  python -c "
import json; d=json.loads(open('$OUT/bench_r02h_$C.json').read().strip().splitlines()[-1])
print('$C', round(d['value']), 'e2e', round(d['e2e']['value'] or 0), 'p50', round(d['latency_ms']['p50'],4), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), d['roofline']['kernel'], round(d['roofline']['frac'],3))
print({k: round(v, 1) for k, v in sorted(d['kernels_us'].items(), key=lambda x: -x[1])})"
done
for P in 1 2; do
  timeout 600 python bench.py --inflight $P --steps 200 --no-cpu-baseline > $OUT/bench_r02h_p$P.json 2> /dev/null
  python -c "
import json; d=json.loads(open('$OUT/bench_r02h_p$P.json').read().strip().splitlines()[-1])
print('c2 P=$P', round(d['value']), 'p50', round(d['latency_ms']['p50'],4), 'p99', round(d['latency_ms']['p99'],4), 'e2e', round(d['e2e']['value']), d['e2e']['ticks_in_flight'])"
done
timeout 600 python bench.py --e2e-inflight 6 --steps 200 --no-cpu-baseline > $OUT/bench_r02h_e6.json 2> /dev/null
python -c "
import json; d=json.loads(open('$OUT/bench_r02h_e6.json').read().strip().splitlines()[-1])
print('c2 e2e P=6', round(d['value']), 'e2e', round(d['e2e']['value']), d['e2e']['ticks_in_flight'], d['e2e']['mode'])"
