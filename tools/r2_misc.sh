set -u
OUT=gpurun_out
bash tools/r2_prof.sh clu line3_cluster --nx 64 --ny 63 --batch 16384
SAN_BATCH=3 SAN_CASES=banded timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_cases.py > $OUT/racecheck_banded_r2.txt 2>&1
echo "rc=$?" >> $OUT/racecheck_banded_r2.txt
SAN_BATCH=3 SAN_CASES=banded timeout 900 compute-sanitizer --tool initcheck python tools/sanitize_cases.py > $OUT/initcheck_banded_r2.txt 2>&1
echo "rc=$?" >> $OUT/initcheck_banded_r2.txt
