# Boltzmann Newton solve: build, GPU parity tests, C2 timing
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_boltzmann.py -m gpu -q -s -x -k "debye or warm or full" > gpurun_out/pytest_boltz1.log 2>&1; tail -15 gpurun_out/pytest_boltz1.log
