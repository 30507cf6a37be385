cp paper_conf_ipps_binderlp19_b200/libsnp_trace.so paper_conf_ipps_binderlp19_b200/libsnp.so
MODE=search timeout 300 python scripts/trace_fastid2.py > gpurun_out/trace2.log 2>&1
MODE=xor timeout 300 python scripts/trace_fastid2.py >> gpurun_out/trace2.log 2>&1
cat gpurun_out/trace2.log
