python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q 2>&1 | grep -vE "^\s*$" | tail -60
