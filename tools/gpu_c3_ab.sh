# C3 HtoD fixed-cost probe on one B200 (tools/c3_htod_ab.py): timings per size and context variant, plus
# serialized launch lists for one 1 MiB and one 64 MiB call.  Outputs under gpurun_out/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
timeout 600 python tools/c3_htod_ab.py ${LOGS:-12,20,22,24,26,28,30} ${VARS:-default,one_cta} > gpurun_out/c3ab.json 2> gpurun_out/c3ab.err
for lg in 20 26; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/c3_launch_$lg.csv \
    python tools/c3_htod_ab.py $lg default > /dev/null 2>&1
done
echo done > gpurun_out/c3ab_done.txt
