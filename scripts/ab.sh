#!/bin/bash
# A/B two builds of libsr.so in one box session: scripts/ab.sh <a.so> <b.so> <reps> <command...>
a=$1; b=$2; n=$3; shift 3
for i in $(seq $n); do
  for v in $a $b; do
    cp $v paper_conf_sigcomm_kimjyyh20_b200/libsr.so
    echo "== $v"; "$@"
  done
done
