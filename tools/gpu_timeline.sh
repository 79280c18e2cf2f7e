#!/bin/bash
# Round-trip per-layer timeline under experiment knobs (which kinds are CUDA-event timed, stream priority)
mkdir -p gpurun_out
run() { n=$1; shift; env "$@" timeout 300 python tools/roundtrip_timeline.py --reps 2 $ARGS > gpurun_out/tl_$n.json 2> gpurun_out/tl_$n.err; }
ARGS="--dma-piece-mib 4096" run fix_timed_all AEG_DEBUG_TIMED_KINDS=15
ARGS="--dma-piece-mib 4096 --no-timing" run fix_untimed AEG_DEBUG_TIMED_KINDS=15
ARGS="--dma-piece-mib 128" run fix_pieces128_timed AEG_DEBUG_TIMED_KINDS=15
