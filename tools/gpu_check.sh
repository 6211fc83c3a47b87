set -x
nvidia-smi -L; free -g | head -2; nproc
python -c "import torch; print(torch.cuda.get_device_name(0))"
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -40 > gpurun_out/pytest_gpu.txt
tail -40 gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
timeout 600 python bench.py --n 268435456 --steps 5 --warmup 3 --no-cpu --e2e-steps 1 2>&1 | tail -5
timeout 900 python bench.py --steps 5 --warmup 3 --cpu-seconds 5 2>&1 | tail -5
