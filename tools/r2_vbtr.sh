#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for o in u64 u256; do for srt in 1 0; do echo "$o sort=$srt"; KAMI_VB_SORT=$srt timeout 300 python tools/trace_vb.py $o 65536 | tail -11; done; done
