for e in 0 128 130 48 176; do echo "== exp $e"; SR_BLOCK_EXP=$e python scripts/bench_block.py 2>&1 | grep -E "^resblock|E1_iss  " | head -8; done
