#!/bin/bash
# one GPU round-trip: device info, build+smoke, parity tests, a short bench (run under gpurun)
mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
python -c "import torch;p=torch.cuda.get_device_properties(0);print(p)"
python -c "import __graft_entry__ as e; e.build(); e.smoke()" 2>&1 | tail -5
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -5
