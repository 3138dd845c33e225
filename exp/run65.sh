python exp/e2e_probe2.py
python exp/e2e_probe.py
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gate.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gate.log
