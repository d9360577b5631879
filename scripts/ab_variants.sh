# A/B several builds of libsr.so (build/ab/<name>.so) in one box session:
#   scripts/ab_variants.sh <reps> <script.py> <names...>   (the script gets the variant name as argv[1])
n=$1; sc=$2; shift 2
for i in $(seq $n); do for v in "$@"; do cp build/ab/$v.so paper_conf_sigcomm_kimjyyh20_b200/libsr.so; python $sc $v; done; done
