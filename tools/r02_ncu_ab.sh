#!/bin/bash
bash tools/ncu_c4max.sh
bash tools/ab_c4max.sh 112 "prio_on||" "prio_off|SH_SIDE_PRIO=0|"
