set -u
OUT=gpurun_out/s3b; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -p no:randomly --timeout 300 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 420 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
VARDIR=varlib KS="6 8 10" bash tools/variant_sweep.sh > $OUT/variants.txt 2>&1
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
cat $OUT/variants.txt
