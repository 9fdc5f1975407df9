# build libsmiler.so variants into _build/var/<name>.so: name=flags pairs
set -e
cd "$(dirname "$0")/.."
mkdir -p paper_conf_sigmod_zhout15_b200/_build/var
for spec in "$@"; do
  name=${spec%%=*}; flags=${spec#*=}
  SMILER_EXTRA_NVFLAGS="$flags" python -c "from paper_conf_sigmod_zhout15_b200.build import build; build(force=True)"
  cp paper_conf_sigmod_zhout15_b200/libsmiler.so paper_conf_sigmod_zhout15_b200/_build/var/$name.so
done
python -c "from paper_conf_sigmod_zhout15_b200.build import build; build(force=True)"
