python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_field.py -x -q 2>&1 | tail -15
timeout 300 python scripts/field_probe.py 2>&1 | tail -25
