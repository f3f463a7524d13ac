#!/bin/bash
# Round 2 (r02c) closing bench lines after the last kernel changes: GPU tests, smoke, C1-C5 and C2 perm,
# C2 launch list.  Outputs gpurun_out/<tag>_*.
set -u
tag=${1:-r02cclose}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${tag}_bench_C3.json 2> gpurun_out/${tag}_bench_C3.err
for c in C1 C2 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/${tag}_bench_$c.json 2> gpurun_out/${tag}_bench_$c.err
done
timeout 300 python bench.py --config C2 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_bench_C2perm.json 2> gpurun_out/${tag}_bench_C2perm.err
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C2.csv python scripts/profile_step.py --config C2 > /dev/null 2>&1
ls gpurun_out | grep $tag
