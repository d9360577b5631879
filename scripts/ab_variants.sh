# A/B several builds of libsr.so (build/ab/<name>.so) in one box session: scripts/ab_variants.sh <reps> <names...>
n=$1; shift
for i in $(seq $n); do for v in "$@"; do cp build/ab/$v.so paper_conf_sigcomm_kimjyyh20_b200/libsr.so; python scripts/bt_time.py $v; done; done
