for c in C5 C3; do for tm in 1 2 4; do echo -n "tau_mult $tm: "; bash tools/bench_brief.sh $c --no-e2e --tau-mult $tm; done; done
