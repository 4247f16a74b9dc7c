# A/B of CTA sizes with per-lane shared arrays sized to the CTA (GSWORD_SMEM_LANES)
set -u
mkdir -p gpurun_out
W=${VB_WORK:-C1:1,C1:2,C1:0,C2:0,C3:0}
VB_WORK=$W python scripts/variant_bench.py build/variants/lib_a_base.so > gpurun_out/abc.jsonl 2> gpurun_out/abc.err
VB_WORK=$W VB_OPTS=1=224 VB_TAG=":t224" python scripts/variant_bench.py build/variants/lib_l_l224.so >> gpurun_out/abc.jsonl 2>> gpurun_out/abc.err
VB_WORK=$W VB_OPTS=1=192 VB_TAG=":t192" python scripts/variant_bench.py build/variants/lib_m_l192.so >> gpurun_out/abc.jsonl 2>> gpurun_out/abc.err
VB_WORK=$W VB_OPTS=1=160 VB_TAG=":t160" python scripts/variant_bench.py build/variants/lib_m_l192.so >> gpurun_out/abc.jsonl 2>> gpurun_out/abc.err
echo done
