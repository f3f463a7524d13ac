#!/bin/bash
# Round-3 measurement suite (GPU box, repo root): GPU tests, smoke, bench lines C1-C5 + reference arm,
# general-CSC (C2 perm) line, launch lists, ncu --set full of the dominant kernels (C3 pre_fused, C4
set -u
tag=${1:-r02cf}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${tag}_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${tag}_bench_C3.json 2> gpurun_out/${tag}_bench_C3.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${tag}_ref.json 2> gpurun_out/${tag}_ref.err
for c in C1 C2 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/${tag}_bench_$c.json 2> gpurun_out/${tag}_bench_$c.err
done
timeout 300 python bench.py --config C2 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_bench_C2perm.json 2> gpurun_out/${tag}_bench_C2perm.err
P="python scripts/profile_step.py"
for c in C3 C4 C5; do
  ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
      --log-file gpurun_out/${tag}_launches_$c.csv $P --config $c > /dev/null 2>&1
done
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C2perm.csv $P --config C2 --mode perm > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:pre_fused --csv --log-file gpurun_out/${tag}_traffic_C3.csv $P --config C3 > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:pre_cluster --csv --log-file gpurun_out/${tag}_traffic_C4.csv $P --config C4 > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:layer_gen --csv --log-file gpurun_out/${tag}_traffic_C2_perm.csv $P --config C2 --mode perm > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_C3 pre_fused 0 1 $P --config C3
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_C4 pre_cluster 0 1 $P --config C4
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen layer_gen 2 1 $P --config C2 --mode perm
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen5 layer_gen 2 1 $P --config C5 --t 18
ls gpurun_out | grep $tag
