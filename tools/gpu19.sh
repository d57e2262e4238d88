python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_kv.py -x -q 2>&1 | tail -30
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
