#!/bin/bash
# Round-2 evidence: bench line, ncu launch list of the bench command, and one ncu --set full
# capture per kernel (bench workloads + tools/prof_extra.py).  Outputs under gpurun_out/r2/.
mkdir -p gpurun_out/r2
export LDDP_TIMEOUT_MS=30000
O=gpurun_out/r2
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c5.csv \
  python bench.py --steps 2 --warmup 3 --no-others --no-cpu > $O/launches_c5.log 2>&1
cap() {   # name, kernel regex, command...
  local name=$1 k=$2; shift 2
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:$k -s ${SKIP:-3} -c 1 \
    -o $O/prof_$name -f "$@" > $O/ncu_$name.log 2>&1
  echo "$name rc=$?" >> $O/caps.txt
}
cap c5_lcs16 lcs16 python bench.py --workload C5 --no-others --no-cpu --steps 1 --warmup 3
cap c1_lcs16 lcs16 python bench.py --workload C1 --no-others --no-cpu --steps 1 --warmup 3
cap c2_adiag adiag python bench.py --workload C2 --no-others --no-cpu --steps 1 --warmup 3
cap c3_fsk fsk python bench.py --workload C3 --no-others --no-cpu --steps 1 --warmup 3
cap c4_prevrow_hx prevrow_hx python bench.py --workload C4 --no-others --no-cpu --steps 1 --warmup 3
cap c6_invl invl python bench.py --workload C6 --no-others --no-cpu --steps 1 --warmup 3
cap c7_prevrow_hx prevrow_hx python bench.py --workload C7 --no-others --no-cpu --steps 1 --warmup 3
cap c8_fsk_batch fsk python bench.py --workload C8 --no-others --no-cpu --steps 1 --warmup 3
SKIP=0 cap x_wavefront_table wavefront python tools/prof_extra.py
SKIP=0 cap x_adiag_table adiag python tools/prof_extra.py
SKIP=0 cap x_traceback traceback python tools/prof_extra.py
SKIP=0 cap x_prevrow_fallback "prevrow_kernel" python tools/prof_extra.py
SKIP=0 cap x_transpose transpose python tools/prof_extra.py
SKIP=0 cap x_invl_mirror invl python tools/prof_extra.py
SKIP=0 cap x_prevrow_cb_table prevrow_cb python tools/prof_extra.py
for f in $O/prof_*.ncu-rep; do
  b=$(basename $f .ncu-rep)
  python tools/ncu_summary.py $f > $O/${b}.json 2>/dev/null
  ncu -i $f --page raw --csv 2>/dev/null | gzip > $O/${b}_raw.csv.gz
done
# keep the two headline reports (C5 lcs16, C4 prevrow_cb); the rest are summarised above
for f in $O/prof_*.ncu-rep; do
  case $f in *c5_lcs16*|*c4_prevrow_hx*) ;; *) rm -f $f ;; esac
done
du -sh $O
