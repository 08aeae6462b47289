#!/bin/bash
# bash tools/knob_sweep.sh > gpurun_out/knob_sweep.txt
cd "$(dirname "$0")/.."
python tools/knob_sweep.py
for b in 4 6 10 12 16; do EGEMM_BAND=$b python tools/knob_sweep.py; done
for pe in 4 16; do EGEMM_PACE_E=$pe python tools/knob_sweep.py; done
for ps in 3 4; do EGEMM_PACE_S=$ps python tools/knob_sweep.py; done
EGEMM_NO_PACE=1 python tools/knob_sweep.py
python tools/knob_sweep.py
