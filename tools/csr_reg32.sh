# a1 rows of <= 32 entries: register bitonic (MP_CSR_REG32=1, default) vs register rank sort (0); parity
# (experiment record: the register bitonic for <= 32-entry rows measured neutral and was removed -- DESIGN "Experiments that did not pay")
set -u
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -1
for rep in 1 2; do for c in c4 c3; do for v in 0 1; do
  echo "== REG32=$v $c"; MP_CSR_REG32=$v timeout 300 python tools/ingest_breakdown.py $c 5 2>&1 | tail -2 | head -1 | python -c "
import sys,ast; l=sys.stdin.read(); d=ast.literal_eval(l[l.index('{'):]); print(l[:l.index('{')], {k:d[k] for k in d if 'rowsort' in k})"
done; done; done
