timeout 300 python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /tmp/b.json 2>/dev/null; echo bench=$?; tail -1 /tmp/b.json | cut -c1-300
