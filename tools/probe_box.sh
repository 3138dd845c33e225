set -x
nvidia-smi
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm,clocks.max.mem --format=csv
nproc; lscpu | head -20; free -g
python - <<'PY'
import torch
p=torch.cuda.get_device_properties(0)
print(p)
print("L2", getattr(p,'L2_cache_size',None), "SMs", p.multi_processor_count, "mem", p.total_memory)
import ctypes
cu=ctypes.CDLL("libcudart.so") if False else None
PY
python -c "import cuda; print('cuda-python ok')"
ncu --version
