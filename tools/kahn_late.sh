# k_kahn: speculative (default) vs late (MP_KAHN_V bit 16) row-range loads, twice each
set -u
for rep in 1 2; do
for c in c3 c4 lu64; do for v in 13 29; do echo "== V=$v $c"; MP_KAHN_V=$v timeout 300 python tools/ingest_breakdown.py $c 5 2>&1 | tail -2 | head -1 | cut -c1-110; done; done
for v in 1 17; do echo "== V=$v c2 colr0"; MP_KAHN_COLR=0 MP_KAHN_V=$v timeout 300 python tools/ingest_breakdown.py c2 5 2>&1 | tail -2 | head -1 | cut -c1-110; done
done
