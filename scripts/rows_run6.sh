export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/rows6; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1; tail -3 $O/tests.log
cd scripts; python small_probe2.py > ../$O/probe.txt 2>&1; cd ..
grep -h "auto dynamic wpc 0 step 0" $O/probe.txt
