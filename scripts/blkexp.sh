for e in 0; do echo "== exp $e"; SR_BLOCK_EXP=$e python scripts/bench_block.py 2>&1 | grep -E "^resblock|E1_iss  " | head -8; done
python -m pytest tests/test_gpu_net.py -q -x 2>&1 | tail -2
