# round-2 evidence after word mode (v23): default bench (C3), C1/C2 lines, reference arm,
# ncu launch list + full capture of the word kernel on C3, sanitizers incl. word mode
bash scripts/gpu_job.sh v23 bench:c3 bench:c1 bench:c2 ncu:c3 sanitize:memcheck sanitize:racecheck sanitize:synccheck
