#!/bin/bash
# Round-end measurement suite (GPU box, repo root): tests, C2 bench + ncu (measure.sh), C1/C3/C4/C5 bench
# lines, C3 ncu capture of the row-resident kernel.  Outputs under gpurun_out/<tag>_*.
set -u
tag=${1:-fin}
mkdir -p gpurun_out
python -m pytest tests -m gpu -q > gpurun_out/${tag}_pytest_gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
scripts/measure.sh ${tag}_C2 C2
for c in C1 C3 C4 C5; do
    python bench.py --config $c > gpurun_out/${tag}_bench_$c.json 2> gpurun_out/${tag}_bench_$c.err
done
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:pre_fused --csv --log-file gpurun_out/${tag}_C3_traffic.csv \
    python scripts/profile_step.py --config C3 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_C3_full pre_fused 0 1 python scripts/profile_step.py --config C3
