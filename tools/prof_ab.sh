#!/bin/bash
# ncu --set full of one launch of workload $W for the shipped library and each
# variant libsb_<name>.so in $LIBS -> gpurun_out/$O/prof_<lib>_$W.ncu-rep
O=gpurun_out/${O:-profab}
mkdir -p $O
W=${W:-C2}
ncu --set full --clock-control none --import-source on -k regex:sb_ -s 2 -c 1 -o $O/prof_main_$W -f \
    python tools/prof_run.py --workload $W --n 3 > $O/prof_main_$W.log 2>&1
for v in $LIBS; do
  SB_LIB_PATH=$PWD/paper_conf_sc_asahilbpbgo24_b200/libsb_$v.so ncu --set full --clock-control none --import-source on \
    -k regex:sb_ -s 2 -c 1 -o $O/prof_${v}_$W -f python tools/prof_run.py --workload $W --n 3 > $O/prof_${v}_$W.log 2>&1
done
ls $O
