# A/B of the k_kahn variants (MP_KAHN_V bits) on the ingest breakdown + build parity tests
set -u
for v in ${VS:-0 1 4 5}; do
  echo "== MP_KAHN_V=$v"
  for c in c2 c3 c4; do MP_KAHN_V=$v timeout 300 python tools/ingest_breakdown.py $c 5 2>&1 | tail -2 | cut -c1-120; done
done
for v in ${TV:-4 5}; do
  MP_KAHN_V=$v timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -2
done
