#!/bin/bash
# Round-2 measurement suite (GPU box, repo root): GPU tests, smoke, default bench + reference arm, ncu launch
# list and --set full captures (C3 dominant kernel, Alg. 2 / residue kernels at C2 t = 10, general CSC),
# FFMA micro-benchmark, compute-sanitizer.  Outputs gpurun_out/<tag>_*.
set -u
tag=${1:-r02f}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${tag}_smi.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q --durations=20 > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${tag}_ref.json 2> gpurun_out/${tag}_ref.err
for c in C1 C2 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/${tag}_bench_$c.json 2> gpurun_out/${tag}_bench_$c.err
done
timeout 300 python scripts/popc_timing.py > gpurun_out/${tag}_popc_C3.txt 2>&1
timeout 300 python scripts/popc_timing.py --config C2 > gpurun_out/${tag}_popc_C2.txt 2>&1
P="python scripts/profile_step.py"
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C3.csv $P --config C3 > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:pre_fused --csv --log-file gpurun_out/${tag}_traffic_C3.csv $P --config C3 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_C3 pre_fused 0 1 $P --config C3
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_res "map_|residual_traj" 0 3 $P --config C2 --t 10
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C2t10.csv $P --config C2 --t 10 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_ell layer_ell 2 1 $P --config C2 --mode perm
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:layer_ell --csv --log-file gpurun_out/${tag}_traffic_C2_perm.csv $P --config C2 --mode perm > /dev/null 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubf scripts/ubench_ffma.cu && /tmp/ubf > gpurun_out/${tag}_ubench_ffma.txt 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python scripts/sanitize.py > gpurun_out/${tag}_sanitizer_$tool.txt 2>&1
done
ls gpurun_out | grep $tag
