#!/bin/bash
# One gpurun session: GPU tests, bench, launch list and ncu captures (outputs in gpurun_out/).
# usage: tools/gpu_session.sh <tag> [tests|bench|ncu ...]
tag=${1:-r01}; shift
what=${@:-tests bench ncu}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${tag}_smi.txt
for w in $what; do
  case $w in
    smoke) timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/${tag}_smoke.log;;
    tests) timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/${tag}_tests.log 2>&1; echo "tests rc=$?";;
    bench) timeout 900 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?"; tail -c 3000 gpurun_out/${tag}_bench.json;;
    benchfast) timeout 600 python bench.py --no-extras > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?"; tail -c 3000 gpurun_out/${tag}_bench.json;;
    ncu)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
        --log-file gpurun_out/${tag}_launches.csv python tools/ncu_target.py --kind acoustic --nt 20 > /dev/null 2>&1; echo "launches rc=$?"
      for k in ac_v ac_p; do
        timeout 600 ncu --set full --clock-control none --import-source on -k regex:${k}_kernel -s 4 -c 1 \
          -o gpurun_out/${tag}_${k} python tools/ncu_target.py --kind acoustic --nt 6 > gpurun_out/${tag}_${k}_ncu.log 2>&1; echo "ncu $k rc=$?"
      done;;
    ncuiso)
      timeout 600 ncu --set full --clock-control none --import-source on -k regex:iso_step -s 2 -c 1 \
        -o gpurun_out/${tag}_iso python tools/ncu_target.py --kind iso --n 512 --nt 4 > gpurun_out/${tag}_iso_ncu.log 2>&1; echo "ncu iso rc=$?";;
    ncuel)
      for k in el_v el_s; do
        timeout 600 ncu --set full --clock-control none --import-source on -k regex:${k}_kernel -s 2 -c 1 \
          -o gpurun_out/${tag}_${k} python tools/ncu_target.py --kind elastic --n 384 --nt 4 > gpurun_out/${tag}_${k}_ncu.log 2>&1; echo "ncu $k rc=$?"
      done;;
  esac
done
