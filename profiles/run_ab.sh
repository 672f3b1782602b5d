# A/B of abvar/ builds against the in-tree library (args: config then variant names)
cfg=$1; shift
bash profiles/ab.sh $cfg "$@" > gpurun_out/ab.txt 2>&1
cat gpurun_out/ab.txt
