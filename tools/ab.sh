# A/B: run "$@" once per library variant in paper_conf_sigmod_zhout15_b200/_build/var/*.so
# (each copied over libsmiler.so in this snapshot), printing the variant name first.
L=paper_conf_sigmod_zhout15_b200/libsmiler.so
cp $L /tmp/libsmiler.base.so
for v in paper_conf_sigmod_zhout15_b200/_build/var/*.so; do
  cp $v $L; echo "== $(basename $v .so)"; "$@"
done
cp /tmp/libsmiler.base.so $L
