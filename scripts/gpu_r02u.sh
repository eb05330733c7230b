#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multigpu.py tests/test_gpu_solvers.py -m gpu -q > gpurun_out/pytest_u.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_u.log
