#!/bin/bash
# Round-2 GPU check (GPU box, repo root): GPU tests (optionally a -k filter), smoke, default bench line.
#   scripts/r02_check.sh <tag> [pytest -k expr]
set -u
tag=$1; kexpr=${2:-}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${tag}_smi.txt 2>&1
nproc >> gpurun_out/${tag}_smi.txt
if [ -n "$kexpr" ]; then
  timeout 1800 python -m pytest tests -m gpu -q -x -k "$kexpr" --durations=15 > gpurun_out/${tag}_pytest_gpu.txt 2>&1
else
  timeout 1800 python -m pytest tests -m gpu -q --durations=25 > gpurun_out/${tag}_pytest_gpu.txt 2>&1
fi
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
echo "bench rc=$?" >> gpurun_out/${tag}_bench.err
