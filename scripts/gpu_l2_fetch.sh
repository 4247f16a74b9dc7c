set -u
mkdir -p gpurun_out
timeout 1200 python scripts/l2_fetch_probe.py -1 32 64 128 > gpurun_out/l2f.jsonl 2> gpurun_out/l2f.err
GRAN=32 timeout 300 ncu --clock-control none -k regex:gather_kernel --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_op_read_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum --csv python -c "
import sys; sys.path.insert(0,'.')
import torch; torch.empty(1,device='cuda')
from cuda.bindings import runtime as rt
print(rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity, 32), rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity))
import paper_journals_pacmmod_yelsg24_b200 as G
with G.Context(0) as ctx:
    for mb in (64, 450, 2048): print(mb, ctx.gather_roofline(mb << 20, 4))
" > gpurun_out/l2f_ncu.csv 2> gpurun_out/l2f_ncu.err
echo done
