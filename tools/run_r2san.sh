timeout 600 python tools/sanitize_target.py 2>&1 | tail -2
bash tools/gpu_sanitize.sh
