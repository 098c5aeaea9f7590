#!/usr/bin/env bash
# One parametrised gpurun job (replaces the round-1 one-off scripts):
#   bash scripts/gpu_job.sh <tag> <step> [<step> ...]
# steps:
#   smoke                  build + __graft_entry__.smoke()
#   pytest[:<expr>]        pytest -m gpu (optionally -k <expr>)
#   bench:<cfg>[:<args>]   bench.py --workload <cfg> (extra args, comma separated)
#   ref[:<cfg>]            bench.py --impl reference
#   ncu:<cfg>[:<cycles>]   launch list + one --set full capture of the dominant kernel
#   sanitize:<tool>        compute-sanitizer <tool> on the short C1/C2 sanitizer run
#   prof:<cfg>             scripts/prof_run.py --phases
# Everything lands in gpurun_out/<tag>_*.
set -u
TAG=$1; shift
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
for s in "$@"; do
  IFS=: read -r kind a b <<< "$s"
  case $kind in
    smoke) timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; tail -1 $O/${TAG}_smoke.log ;;
    pytest) if [ -n "$a" ]; then K=(-k "$a"); else K=(); fi
            timeout 2400 python -m pytest tests -m gpu -x -q "${K[@]}" > $O/${TAG}_pytest.log 2>&1; tail -3 $O/${TAG}_pytest.log ;;
    bench) X=${b//,/ }
           timeout 900 python bench.py --workload $a $X > $O/${TAG}_bench_$a.json 2> $O/${TAG}_bench_$a.err
           tail -c 400 $O/${TAG}_bench_$a.json; tail -3 $O/${TAG}_bench_$a.err ;;
    ref) timeout 900 python bench.py --impl reference --workload ${a:-c3} > $O/${TAG}_ref_${a:-c3}.json 2> $O/${TAG}_ref.err; tail -c 300 $O/${TAG}_ref_${a:-c3}.json ;;
    ncu) C=${b:-0}; [ "$C" = 0 ] && C=$(python -c "print({'c4':200,'c5':100}.get('$a',1000))")
         timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_$a.csv \
           python bench.py --workload $a --steps 2 --warmup 3 --cycles $C --no-cpu-baseline --no-batched > /dev/null 2>&1
         K=$(python -c "print('gem_lane_kernel' if '$a'=='c5' else 'gem_(step|word)_kernel')")
         timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:$K" -s 1 -c 1 -f -o $O/${TAG}_ncu_$a \
           python scripts/prof_run.py --cfg $a --cycles $C --streams $( [ "$a" = c5 ] && echo 4096 || echo 1 ) > /dev/null 2>&1
         python scripts/ncu_summary.py $O/${TAG}_launches_$a.csv $O/${TAG}_ncu_$a.ncu-rep $O/${TAG}_ncu_$a $C > /dev/null 2>&1
         head -12 $O/${TAG}_ncu_$a.md ;;
    sanitize) timeout 1500 compute-sanitizer --tool $a --error-exitcode 9 python scripts/sanitize_run.py > $O/${TAG}_sanitize_$a.log 2>&1
              echo "sanitize $a rc=$?"; tail -5 $O/${TAG}_sanitize_$a.log ;;
    prof) timeout 600 python scripts/prof_run.py --cfg $a --phases > $O/${TAG}_prof_$a.log 2>&1; tail -8 $O/${TAG}_prof_$a.log ;;
    *) echo "unknown step $s" ;;
  esac
done
