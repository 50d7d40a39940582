./scripts/micro/gridsync
timeout 300 python scripts/field_probe.py 2>&1 | tail -12
