timeout 600 python -m pytest tests/test_gpu_field.py tests/test_gpu_multirank.py -x -q 2>&1 | tail -15
