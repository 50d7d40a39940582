python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python scripts/debug_mr4.py 2>&1 | tail -8
timeout 600 python scripts/debug_mr3.py 2>&1 | head -2
OPP_REFILL=1 timeout 600 python scripts/debug_mr3.py 2>&1 | head -1
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3
