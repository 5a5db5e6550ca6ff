#!/bin/bash
T=${1:-r2i}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -k "detail" -m gpu -q -rf --tb=short --timeout 240 > gpurun_out/${T}_detail.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_detail.log
bash tools/gpu_evidence_r2.sh ev2
