# lcs16: group-unroll sweep + one ncu capture of C5 (development script)
mkdir -p gpurun_out
for GU in 1 2 4; do
LDDP_L16_GU=$GU timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --no-others --no-cpu > gpurun_out/l16_gu$GU.json 2>&1
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:lcs16 -s 2 -c 1 -o gpurun_out/prof_l16_C5 -f python bench.py --workload C5 --steps 1 --warmup 3 --no-others --no-cpu > gpurun_out/ncu_l16.log 2>&1
