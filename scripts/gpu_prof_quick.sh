set -u
mkdir -p gpurun_out
make all > gpurun_out/p_build.log 2>&1
python -c "
import torch
p=torch.cuda.get_device_properties(0); print(p)
from cuda.bindings import runtime as rt
for a in ('cudaDevAttrMaxPersistingL2CacheSize','cudaDevAttrMaxAccessPolicyWindowSize','cudaDevAttrL2CacheSize'):
    print(a, rt.cudaDeviceGetAttribute(getattr(rt.cudaDeviceAttr,a),0))
" > gpurun_out/p_attrs.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:sample_kernel -c 2 \
    -o gpurun_out/p_full python scripts/profile_driver.py --samples 1e8 --l2 2 > gpurun_out/p_full.log 2>&1
python scripts/ncu_lines.py gpurun_out/p_full.ncu-rep "" 60 > gpurun_out/p_lines.txt 2>&1
ls -la gpurun_out
