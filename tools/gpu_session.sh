#!/bin/bash
# One gpurun session: GPU test suite, probe-build diagnostics, bench.
#   gpurun --timeout 2400 -- 'bash tools/gpu_session.sh <tag> [what...]'
# what: tests | suitor | parts | bench | ncu_<kernel-regex>   (default: tests parts bench)
TAG=${1:-run}; shift
WHAT=${@:-tests parts bench}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt 2>&1
lscpu | grep -E "Model name|^CPU\(s\)" > $OUT/host.txt 2>&1; free -g >> $OUT/host.txt 2>&1
PROBES=$PWD/paper_conf_sc_xiangkfah23_b200/lib/libcualign_bp_probes.so
for w in $WHAT; do
  case $w in
    tests)
      timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=15 > $OUT/pytest.txt 2>&1
      echo "pytest rc=$?"; tail -25 $OUT/pytest.txt ;;
    suitor)
      CUALIGN_LIB=$PROBES CUALIGN_MATCH_DEBUG=1 timeout 300 python tools/probe_suitor.py > $OUT/suitor.txt 2>&1
      echo "suitor rc=$?"; tail -20 $OUT/suitor.txt ;;
    parts)
      timeout 300 python tools/bench_parts.py --pre 80 --n 50 > $OUT/parts.json 2> $OUT/parts.err
      echo "parts rc=$?"; cat $OUT/parts.json ;;
    pp_*)
      # parts with the probe build and env assignments: pp_NAME=VAL,NAME2=VAL2
      ENVS=$(echo ${w#pp_} | tr ',' ' ')
      env CUALIGN_LIB=$PROBES $ENVS timeout 300 python tools/bench_parts.py --pre 80 --n 50 > $OUT/parts_${w}.json 2> $OUT/parts_${w}.err
      echo "$w rc=$?"; cat $OUT/parts_${w}.json ;;
    shardtests)
      timeout 900 python -m pytest tests/test_gpu_shard.py tests/test_gpu_nccl.py tests/test_gpu_layout.py -q -p no:cacheprovider > $OUT/shardtests.txt 2>&1
      echo "shardtests rc=$?"; tail -5 $OUT/shardtests.txt ;;
    n2)
      bash tools/run_bench_n2_onegpu.sh $TAG ;;
    knntests)
      timeout 600 python -m pytest tests/test_gpu_knn.py -q -p no:cacheprovider > $OUT/knntests.txt 2>&1
      echo "knntests rc=$?"; tail -3 $OUT/knntests.txt ;;
    knn_*)
      ENVS=$(echo ${w#knn_} | tr ',' ' ')
      env CUALIGN_LIB=$PROBES $ENVS timeout 600 python tools/bench_knn.py > $OUT/$w.jsonl 2> $OUT/$w.err
      echo "$w rc=$?"; cat $OUT/$w.jsonl ;;
    sched)
      timeout 1200 python tools/probe_schedules.py > $OUT/sched.jsonl 2> $OUT/sched.err
      echo "sched rc=$?"; cat $OUT/sched.jsonl ;;
    sched_*)
      # schedule probe on O with the probe build and env: sched_NAME=V,NAME2=V
      ENVS=$(echo ${w#sched_} | tr ',' ' ')
      env CUALIGN_LIB=$PROBES $ENVS timeout 600 python tools/probe_schedules.py --points O > $OUT/$w.jsonl 2> $OUT/$w.err
      echo "$w rc=$?"; cat $OUT/$w.jsonl ;;
    steps)
      timeout 600 python tools/probe_steps.py > $OUT/steps.json 2> $OUT/steps.err
      echo "steps rc=$?"; python -c "
import json; d=json.load(open('$OUT/steps.json')); ms=d['ms_per_step']
print('ms per step, first 40:', ms[:40]); print('mean 6-25', sum(ms[5:25])/20, 'mean 60-120', sum(ms[60:])/len(ms[60:]))
[print(x) for x in d['split']]" ;;
    driver)
      # what the driver runs at round end (1 GPU): smoke, bench (20/5), reference arm
      ( time python -c "import __graft_entry__ as g; g.smoke()" ) > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -4 $OUT/smoke.txt
      ( time timeout 1700 python bench.py --gpus 1 --steps 20 --warmup 5 ) > $OUT/bench_driver.json 2> $OUT/bench_driver.err; echo "bench rc=$?"; tail -4 $OUT/bench_driver.err; head -c 600 $OUT/bench_driver.json
      ( time timeout 1700 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 ) > $OUT/ref_driver.json 2> $OUT/ref_driver.err; echo "ref rc=$?"; tail -4 $OUT/ref_driver.err; head -c 400 $OUT/ref_driver.json ;;
    bench)
      timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err
      echo "bench rc=$?"; cut -c1-1500 $OUT/bench.json ;;
    sanitize)
      for tool in memcheck racecheck synccheck initcheck; do
        timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_workload.py > $OUT/sanitize_$tool.txt 2>&1
        echo "sanitize $tool rc=$?"; tail -4 $OUT/sanitize_$tool.txt
      done ;;
    bs_*)
      # the driver's bench window with a forced step schedule (product build): bs_1 pipelined, bs_2 serial, bs_3 forked
      timeout 600 python bench.py --schedule ${w#bs_} --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/$w.json 2> $OUT/$w.err
      timeout 600 python bench.py --schedule ${w#bs_} --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/${w}_300.json 2> $OUT/${w}_300.err
      echo "$w rc=$?"; python -c "
import json
for f in ('$OUT/$w.json', '$OUT/${w}_300.json'):
    d = json.load(open(f)); print(f, round(d['value'],1), {k: round(v,4) for k,v in d['kernel_ms_per_step'].items()})" ;;
    bw_*)
      # the driver's bench window (20 steps after 5) with the probe build and env: bw_NAME=V,NAME2=V
      ENVS=$(echo ${w#bw_} | tr ',' ' ')
      env CUALIGN_LIB=$PROBES $ENVS timeout 600 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/$w.json 2> $OUT/$w.err
      echo "$w rc=$?"; python -c "import json; d=json.load(open('$OUT/$w.json')); print(round(d['value'],1), {k: round(v,4) for k,v in d['kernel_ms_per_step'].items()})" ;;
    initp)
      # init phase trace (probe build), first and later handles
      CUALIGN_LIB=$PROBES CUALIGN_INIT_TRACE=1 timeout 300 python tools/probe_init.py O > $OUT/initp.txt 2>&1
      echo "initp rc=$?"; cat $OUT/initp.txt | tail -40 ;;
    fp32)
      # NEXT-3: fp32 S^p storage, driver window and 300 steps
      timeout 600 python bench.py --fp32 --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/fp32_w.json 2> $OUT/fp32_w.err
      timeout 600 python bench.py --fp32 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/fp32.json 2> $OUT/fp32.err
      echo "fp32 rc=$?"; python -c "
import json
for f in ('$OUT/fp32_w.json', '$OUT/fp32.json'):
    d = json.load(open(f)); print(f, round(d['value'], 1), d['roofline'], d['kernels_isolated']['square'])" ;;
    timeline)
      timeout 300 python tools/probe_timeline.py --pre 10 --n 3 > $OUT/timeline.json 2> $OUT/timeline.err
      echo "timeline rc=$?"; python -c "
import json; d=json.load(open('$OUT/timeline.json'))
for k in d['kernels']: print(k['t0_us'], k['t1_us'], k['dur_us'], k['stream'], k['kernel'])" ;;
    kernw)
      # in-situ per-kernel durations inside the driver's window (p = 6 .. 25)
      timeout 300 python tools/probe_kernels.py --pre 5 --n 20 > $OUT/kernw.json 2> $OUT/kernw.err
      echo "kernw rc=$?"; python -c "import json,sys; d=json.load(open('$OUT/kernw.json')); [print(p, {k: round(v['us_per_step'],1) for k,v in d[p].items()}) for p in d]" ;;
    kern*)
      # in-situ per-kernel durations (CUPTI via torch.profiler); kern or kern_ENV=V,ENV2=V
      ENVS=""; LIBENV=""
      if [ "$w" != "kern" ]; then ENVS=$(echo ${w#kern_} | tr ',' ' '); LIBENV="CUALIGN_LIB=$PROBES"; fi
      env $LIBENV $ENVS timeout 300 python tools/probe_kernels.py --pre 80 --n 20 > $OUT/$w.json 2> $OUT/$w.err
      echo "$w rc=$?"; python -c "import json,sys; d=json.load(open('$OUT/$w.json')); [print(p, {k: round(v['us_per_step'],1) for k,v in d[p].items()}) for p in d]" ;;
    launchlist)
      # the bench command's launch list (cold-cache, serialised: compare shares)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches_bench.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/launchlist.log 2>&1
      echo "launchlist rc=$?"; python tools/launches.py $OUT/launches_bench.csv | head -25 ;;
    ncufp32)
      timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_square_tma -s 10 -c 1 -o $OUT/ncu_sq32 -f python bench.py --fp32 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/ncu_sq32.log 2>&1
      echo "ncufp32 rc=$?"; tail -2 $OUT/ncu_sq32.log ;;
    nculist)
      # launch list (cold-cache, serialised) of a round-only replay at a fixed state
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_propose|k_suitor|k_collect|k_eval|k_mate" -s 100 -c 60 --csv --log-file $OUT/launches_round.csv python tools/bench_parts.py --pre 80 --n 20 > $OUT/nculist.log 2>&1
      echo "nculist rc=$?"; python tools/launches.py $OUT/launches_round.csv 2>/dev/null | head -20 ;;
    ncuparts_*)
      K=${w#ncuparts_}
      timeout 900 ncu --set full --import-source on --clock-control none -k regex:$K -s 20 -c 1 -o $OUT/ncu_$K -f python tools/bench_parts.py --pre 80 --n 10 > $OUT/ncu_$K.log 2>&1
      echo "ncu $K rc=$?"; tail -2 $OUT/ncu_$K.log ;;
    ncu_*)
      K=${w#ncu_}
      timeout 900 ncu --set full --import-source on --clock-control none -k regex:$K -s 10 -c 1 -o $OUT/ncu_$K -f python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-knn --no-configs > $OUT/ncu_$K.log 2>&1
      echo "ncu $K rc=$?"; tail -3 $OUT/ncu_$K.log ;;
  esac
done
