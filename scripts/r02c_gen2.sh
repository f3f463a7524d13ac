#!/bin/bash
set -u
tag=${1:-r02cm}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_round2c.py tests/test_gpu_parity.py -q -x -k "gen or ell or perm or medium or ragged or random or uncompressed or post_modes or c1_vs or pre_fused" > gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest.txt
timeout 300 python bench.py --config C5 --quick --no-cpu-baseline > gpurun_out/${tag}_C5.json 2> gpurun_out/${tag}_C5.err
timeout 300 python bench.py --config C5 --t 18 --quick --no-cpu-baseline > gpurun_out/${tag}_C5u.json 2> gpurun_out/${tag}_C5u.err
timeout 300 python bench.py --config C1 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_C1perm.json 2> gpurun_out/${tag}_C1perm.err
timeout 300 python bench.py --config C2 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_C2perm.json 2> gpurun_out/${tag}_C2perm.err
P="python scripts/profile_step.py"
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen5 layer_gen 2 1 $P --config C5 --t 18
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C5t8.csv $P --config C5 --t 8 > /dev/null 2>&1
ls gpurun_out | grep $tag
