mkdir -p gpurun_out
LDDP_DEBUG=2 timeout 600 ncu --set full --import-source on --clock-control none -k regex:lcs16 -s 2 -c 1 -o gpurun_out/prof_l16_nohand -f python bench.py --workload C5 --steps 1 --warmup 3 --no-others --no-cpu > gpurun_out/ncu_l16n.log 2>&1
