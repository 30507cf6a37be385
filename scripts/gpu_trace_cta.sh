bash scripts/gpu_ab.sh dyn4 libsnp_headA.so libsnp.so libsnp_nodyn.so | cut -c1-170
SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_prof.so timeout 300 python scripts/trace_cta.py
