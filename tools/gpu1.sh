set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -20
timeout 1200 python -m pytest tests -m gpu -x -q -k "not one_epoch" 2>&1 | tail -40
