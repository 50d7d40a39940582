python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python scripts/debug_mr4.py 2>&1 | tail -8
for tg in 1 64; do OPP_TILE_GROUP=$tg timeout 600 python scripts/debug_mr3.py 2>&1 | head -1; done
