python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 python scripts/debug_mr.py 2>&1 | tail -12
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q 2>&1 | grep -E "Error|assert|^E " | head -20
