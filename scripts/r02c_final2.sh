#!/bin/bash
# Round 2 (r02c) closing measurements after R34: GPU tests, smoke, C3 / C2 / C1 bench lines, C3 launch list,
# DRAM traffic and ncu --set full of the dominant kernel.  Outputs gpurun_out/<tag>_*.
set -u
tag=${1:-r02cfin}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${tag}_bench_C3.json 2> gpurun_out/${tag}_bench_C3.err
for c in C1 C2; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/${tag}_bench_$c.json 2> gpurun_out/${tag}_bench_$c.err
done
P="python scripts/profile_step.py"
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C3.csv $P --config C3 > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:pre_fused --csv --log-file gpurun_out/${tag}_traffic_C3.csv $P --config C3 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_C3 pre_fused 0 1 $P --config C3
ls gpurun_out | grep $tag
