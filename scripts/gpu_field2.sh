timeout 600 python -m pytest tests/test_gpu_field.py -x -q 2>&1 | tail -3
timeout 300 python scripts/field_probe.py 2>&1 | tail -25
