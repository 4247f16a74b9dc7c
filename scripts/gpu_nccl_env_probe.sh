mkdir -p gpurun_out
env | grep -i nccl > gpurun_out/envp.txt
python -c "
import os,torch,torch.distributed as dist
os.environ.setdefault('MASTER_ADDR','127.0.0.1'); os.environ.setdefault('MASTER_PORT','29533')
torch.cuda.set_device(0)
dist.init_process_group('nccl', rank=0, world_size=1, device_id=torch.device('cuda',0))
t=torch.ones(4,device='cuda'); dist.all_reduce(t); torch.cuda.synchronize(); print('JSON')
dist.destroy_process_group()
" > gpurun_out/envp_default.out 2> gpurun_out/envp_default.err
NCCL_DEBUG_FILE=/dev/stderr python -c "
import os,torch,torch.distributed as dist
os.environ.setdefault('MASTER_ADDR','127.0.0.1'); os.environ.setdefault('MASTER_PORT','29534')
torch.cuda.set_device(0)
dist.init_process_group('nccl', rank=0, world_size=1, device_id=torch.device('cuda',0))
t=torch.ones(4,device='cuda'); dist.all_reduce(t); torch.cuda.synchronize(); print('JSON')
dist.destroy_process_group()
" > gpurun_out/envp_file.out 2> gpurun_out/envp_file.err
echo done
