python -c "import __graft_entry__ as g; g.build()"
timeout 600 python bench.py --steps 5 --warmup 3 2>&1 | tail -3
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 2>&1 | tail -2
