C="16384,1024,4096,bias_resid 16384,1024,1024,bias_resid 16384,3072,1024,bias 16384,4096,1024,bias_gelu 50432,768,3072,bias_resid 50432,2304,768,bias 50432,3072,768,bias_gelu"
for bn in 0 256 128; do echo "BN=$bn"; E3_GEMM_BN=$bn python scripts/gemm_sweep.py $C; done
