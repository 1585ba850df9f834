set -x
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc" 2>&1 | tail -2
bash scripts/gpu_ssdc_ncu.sh
