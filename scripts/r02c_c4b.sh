#!/bin/bash
set -u
tag=${1:-r02ck}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py -q -x -k "pre_fused or range or cluster" > gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest.txt
timeout 400 python bench.py --config C4 --quick --no-cpu-baseline --pre-fused 4 > gpurun_out/${tag}_C4pf4.json 2> gpurun_out/${tag}_C4pf4.err
timeout 300 python bench.py --config C3 --quick --no-cpu-baseline --pre-fused 4 > gpurun_out/${tag}_C3pf4.json 2> gpurun_out/${tag}_C3pf4.err
ls gpurun_out | grep $tag
