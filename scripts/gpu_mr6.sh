python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for i in 1 2 3 4 5; do timeout 300 python -m pytest tests/test_gpu_multirank.py -q -x 2>&1 | tail -1; done
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_multirank.py -q -x -k "0-2" 2>&1 | grep -vE "^\s*$" | head -60
