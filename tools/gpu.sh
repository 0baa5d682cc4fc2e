#!/bin/bash
# One parametrised recipe for the GPU box (replaces the round-1 one-off
# tools/gpu_run*.sh scripts).  Run through gpurun from the repo root, e.g.
#   gpurun --timeout 1200 -- 'bash tools/gpu.sh TAG tests bench ncu:"--config 5 --m 32 --n 32 --score-bits 7"'
# Every artefact lands in gpurun_out/TAG_*.  Steps (in the order given):
#   tests            pytest -m gpu (junit + log)
#   smoke            __graft_entry__.smoke()
#   bench[:ARGS]     python bench.py ARGS (default: the driver's N=1 command)
#   launches[:ARGS]  ncu launch list (gpu__time_duration, clocks not locked) of bench.py ARGS
#   ncu[:ARGS]       ncu --set full --import-source of the first sweep launch of bench.py ARGS
#                    (exported to TAG_fullI_raw.csv + TAG_fullI_src.csv.gz; KEEP_REP=1 keeps the .ncu-rep)
#   ncupack[:ARGS]   the same for the first pack_kernel launch
#   sanitize         compute-sanitizer memcheck/racecheck/synccheck/initcheck over tests/sanitize_run.py
#   py:FILE[:ARGS]   python FILE ARGS
#   sh:CMD           bash -c CMD (output in TAG_shI.log)
set -u
tag=$1; shift
out=gpurun_out
mkdir -p $out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > $out/${tag}_gpu.txt 2>&1
i=0
for step in "$@"; do
  i=$((i + 1))
  kind=${step%%:*}
  args=""
  [ "$kind" != "$step" ] && args=${step#*:}
  echo "== [$i] $kind $args" | tee -a $out/${tag}_steps.log
  case $kind in
    tests) timeout 1500 python -m pytest tests -m gpu -q --junitxml=$out/${tag}_junit.xml > $out/${tag}_tests.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log ;;
    smoke) timeout 600 python -c 'import __graft_entry__ as g; g.smoke()' > $out/${tag}_smoke.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log ;;
    bench) timeout 1800 python bench.py $args > $out/${tag}_bench$i.json 2> $out/${tag}_bench$i.err; echo "rc=$?" >> $out/${tag}_steps.log ;;
    launches) timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $out/${tag}_launches$i.csv python bench.py $args > $out/${tag}_launches$i.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log ;;
    # ncu full capture of the first sweep launch; the report is exported to
    # text (raw metrics csv + gzipped per-SASS source counters) and deleted
    # unless KEEP_REP=1 (gpurun copies back at most 64 MiB)
    ncu|ncupack) kre=sw_sweep; [ "$kind" = ncupack ] && kre=pack_kernel
       timeout 1800 ncu --set full --clock-control none --import-source on -k regex:$kre -c 1 -o $out/${tag}_full$i python bench.py $args > $out/${tag}_ncu$i.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log
       ncu -i $out/${tag}_full$i.ncu-rep --page raw --csv > $out/${tag}_full${i}_raw.csv 2>/dev/null
       ncu -i $out/${tag}_full$i.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > $out/${tag}_full${i}_src.csv.gz
       [ "${KEEP_REP:-0}" = 1 ] || rm -f $out/${tag}_full$i.ncu-rep ;;
    sanitize) for tool in memcheck racecheck synccheck initcheck; do timeout 1200 compute-sanitizer --tool $tool python tests/sanitize_run.py > $out/${tag}_san_$tool.log 2>&1; echo "$tool rc=$?" >> $out/${tag}_steps.log; done ;;
    py) f=${args%%:*}; a=""; [ "$f" != "$args" ] && a=${args#*:}; timeout 2400 python $f $a > $out/${tag}_py$i.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log ;;
    sh) timeout 2400 bash -c "$args" > $out/${tag}_sh$i.log 2>&1; echo "rc=$?" >> $out/${tag}_steps.log ;;
    *) echo "unknown step $kind" >> $out/${tag}_steps.log ;;
  esac
done
echo done >> $out/${tag}_steps.log
