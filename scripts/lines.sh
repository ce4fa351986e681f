#!/bin/bash
# usage: scripts/lines.sh <rep> [N] [fn-regex]  -- per-source-line attribution for k_gather<VALS=1,SpmvEpi>
rep=$1; n=${2:-40}; fn=${3:-_ZN3inl8k_gatherILb1ENS_7SpmvEpiEEEvNS_10GatherPlanENS_10GatherArgsET0_}
d=$(mktemp -d); (cd $d && cuobjdump -xelf all /root/repo/paper_conf_icpp_liwb15_b200/libinl.so > /dev/null)
cub=$d/spmv.sm_100a.cubin
python /root/repo/scripts/ncu_lines.py $rep ${CUBIN:-$cub} $fn $n
rm -rf $d
