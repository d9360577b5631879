#!/bin/bash
# usage: scripts/prof.sh <out-name> <kernel-regex> <skip> <count> -- <command...>
out=$1; kre=$2; skip=$3; cnt=$4; shift 5
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$kre" -s $skip -c $cnt -o gpurun_out/$out "$@"
