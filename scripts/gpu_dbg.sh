python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 python scripts/debug_tiled.py 2>&1 | tail -20
