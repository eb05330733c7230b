nproc; free -g | head -2; lscpu | grep -E "Model name|Socket|Thread|Core"; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv
python -c "
import torch
p=torch.cuda.get_device_properties(0)
print(p)
print('L2', p.L2_cache_size if hasattr(p,'L2_cache_size') else None)
"
ncu --query-metrics --chip gb100 2>/dev/null | grep -E "^(dram__bytes|lts__t_sector_hit|sm__pipe_fp64|sm__pipe_tensor|sm__inst_executed_pipe_fp64|sm__pipe_fma|sm__inst_executed_pipe_tensor|l1tex__t_requests|l1tex__data_pipe)" | head -60
