set -u
mkdir -p gpurun_out
python scripts/gather_ncu.py > gpurun_out/gn_plain.log 2>&1
timeout 600 ncu --clock-control none -k regex:gather_kernel --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_op_read_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum --csv python scripts/gather_ncu.py > gpurun_out/gn_ncu.csv 2> gpurun_out/gn_ncu.err
timeout 900 ncu --clock-control none --profile-from-start off -k regex:sample_kernel -c 2 --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_op_read_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,lts__t_sectors_srcunit_tex_aperture_device_op_read_lookup_miss.sum --csv python scripts/profile_driver.py --samples 1e8 --l2 2 > gpurun_out/gn_alley.csv 2> gpurun_out/gn_alley.err
echo done
