#!/bin/bash
# Usage (on the GPU box): scripts/ncu_capture.sh <name> <kernel-regex> <skip> <count> <command...>
# One `ncu --set full` capture; the report stays in /tmp, CSV pages (raw, details, SASS source) go to
# gpurun_out/<name>.*.csv (the .ncu-rep itself is too large to bring back).
set -u
name=$1; kre=$2; skip=$3; cnt=$4; shift 4
mkdir -p /tmp/ncu gpurun_out
ncu --set full --clock-control none --import-source on ${NCU_EXTRA:-} -k "regex:$kre" -s "$skip" -c "$cnt" -f -o /tmp/ncu/$name "$@" > gpurun_out/$name.log 2>&1
ncu -i /tmp/ncu/$name.ncu-rep --page raw --csv > gpurun_out/$name.raw.csv
ncu -i /tmp/ncu/$name.ncu-rep --page details --csv > gpurun_out/$name.details.csv
ncu -i /tmp/ncu/$name.ncu-rep --page source --csv --print-source sass > gpurun_out/$name.src.csv 2>/dev/null
