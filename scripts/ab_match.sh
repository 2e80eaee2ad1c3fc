set -u
OUT=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/ -q -x -m gpu 2>&1 | tail -2
for C in c3 c2 c1; do
  for LN in ${LANES:-0}; do
    timeout 600 python bench.py --config $C --steps 100 --warmup 5 --no-cpu-baseline --match-lanes $LN > $OUT/m_${LN}_$C.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/m_${LN}_$C.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('lanes=$LN $C', round(d['value']), 'steady', round(d.get('steady_state',{}).get('value',0) if isinstance(d.get('steady_state'),dict) else 0), {n: round(v,1) for n,v in k.items() if 'match' in n or 'window' in n})"
  done
done
