#!/bin/bash
# The GPU suite against a BZK_CHECK build (device-side bounds asserts; compute-sanitizer is closed on the
# pool), then the new knob tests against the product build
TAG=${1:-r02chk}
mkdir -p gpurun_out
BZK_LIB=$PWD/paper_conf_asplos_lucw0cz25_b200/libbzk_chk.so timeout 2400 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_chk_$TAG.log 2>&1; echo "pytest chk rc=$?"; tail -3 gpurun_out/pytest_gpu_chk_$TAG.log
timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_multiround.py -q > gpurun_out/pytest_knobs_$TAG.log 2>&1; echo "pytest knobs rc=$?"; tail -3 gpurun_out/pytest_knobs_$TAG.log
