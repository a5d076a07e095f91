# A/B of multi-step CUDA graphs (CLOVER_GRAPH_STEPS; variants built by
# scripts/ab_variants.py base= g2=CLOVER_GRAPH_STEPS=2 g4=... g5=... g8=...)
for v in g8 g5; do CLOVER_LIB=build_ab/libclover_$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "graphs or bm64 or tiny or c2_960 or full_size" 2>&1 | tail -1; done
for i in 1 2; do python scripts/ab_variants.py --run base= g2= g4= g5= g8=; done
