bash tools/gpu_ncu_r2.sh r2b
bash tools/gpu_sanitize.sh r2b_san
