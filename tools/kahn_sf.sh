# k_kahn: shared-memory frontier (one block) + speculative row_ptr loads -- parity and A/B
set -u
mkdir -p gpurun_out/ks
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/ks/parity.log 2>&1; echo parity=$?; tail -2 gpurun_out/ks/parity.log
for sf in 0 1; do
  for c in c2 c3 c4; do echo "== SF=$sf $c"; MP_KAHN_SF=$sf timeout 300 python tools/ingest_breakdown.py $c 5 2>&1 | tail -2 | cut -c1-160; done
done
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/ks/bench_c5.json 2> gpurun_out/ks/bench_c5.err; echo c5=$?
python -c "import json;d=json.loads(open('gpurun_out/ks/bench_c5.json').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['roofline']['per_kernel_ms_per_step'])"
