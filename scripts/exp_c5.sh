#!/bin/bash
# C5 global sweep mapping sweep vs the 2R:1W HBM ceiling (scripts/peak_mix.py: torch add 7.10 TB/s)
b() { echo -n "$1: "; shift; env "$@" bash scripts/bench_brief.sh C5 --no-e2e --steps 10; }
b default X=1
b pingpong0 ASTITCH_PINGPONG=0
b U2 ASTITCH_FORCE_UNROLL=2
b U8 ASTITCH_FORCE_UNROLL=8
b thr1024 ASTITCH_FORCE_THREADS=1024
b thr1024_U2 ASTITCH_FORCE_THREADS=1024 ASTITCH_FORCE_UNROLL=2
b thr256_bps2 ASTITCH_FORCE_THREADS=256 ASTITCH_FORCE_BPS=2
b thr256_bps3_U2 ASTITCH_FORCE_THREADS=256 ASTITCH_FORCE_BPS=3 ASTITCH_FORCE_UNROLL=2
b bps2_U2 ASTITCH_FORCE_BPS=2 ASTITCH_FORCE_UNROLL=2
b st_cs ASTITCH_ST_HINT=.cs
