#!/bin/bash
# Round 2 (r02c): general-CSC kernel check (GPU box, repo root).  Outputs gpurun_out/<tag>_*.
set -u
tag=${1:-r02cg}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_round2c.py tests/test_gpu_parity.py -q -x -k "gen or ell or perm or medium or ragged or random or uncompressed or post_modes" > gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest.txt
for g in 1 0; do
  SNICIT_GEN=$g timeout 300 python bench.py --config C2 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_C2perm_gen$g.json 2> gpurun_out/${tag}_C2perm_gen$g.err
  SNICIT_GEN=$g timeout 300 python bench.py --config C5 --t 18 --quick --no-cpu-baseline > gpurun_out/${tag}_C5u_gen$g.json 2> gpurun_out/${tag}_C5u_gen$g.err
done
SNICIT_GEN=1 timeout 300 python bench.py --config C1 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_C1perm_gen1.json 2> gpurun_out/${tag}_C1perm_gen1.err
SNICIT_GEN=1 timeout 300 python bench.py --config C5 --quick --no-cpu-baseline > gpurun_out/${tag}_C5_gen1.json 2> gpurun_out/${tag}_C5_gen1.err
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen layer_gen 2 1 python scripts/profile_step.py --config C2 --mode perm
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen5 layer_gen 2 1 python scripts/profile_step.py --config C5 --t 18 --kernel ell
ls gpurun_out | grep $tag
