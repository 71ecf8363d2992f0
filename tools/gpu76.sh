timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -1
bash tools/gpu65.sh
