bash scripts/gpu_final3.sh
VARS="base5 tminb12 tminb6" bash scripts/gpu_variants.sh
