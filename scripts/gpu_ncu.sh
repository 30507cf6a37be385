# one ncu --set full capture of the top kernel of a workload: WL, KREGEX, SKIP env
set -x
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-tc4_kernel} -s ${SKIP:-4} -c 1 -o gpurun_out/prof_${WL:-fastid1m} python bench.py --workload ${WL:-fastid1m} --steps 2 --warmup 3 --variant ${VAR:-tc} --no-cpu-baseline --no-e2e > gpurun_out/ncu_${WL:-fastid1m}.log 2>&1; echo ncu=$?
