python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 300 python scripts/debug_mr2.py 3 0 2>&1 | tail -20
timeout 300 python scripts/debug_mr2.py 3 2 2>&1 | tail -20
