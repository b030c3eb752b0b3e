# build the working tree → lib/libastra.so, and HEAD's version of the given files → lib/libastra_base.so
set -e
cd /root/repo
python paper_conf_asplos_sivathanucsz19_b200/build.py > /dev/null
cp paper_conf_asplos_sivathanucsz19_b200/lib/libastra.so /tmp/libastra_new.so
git stash push -q -- "$@"
python paper_conf_asplos_sivathanucsz19_b200/build.py > /dev/null || true
cp paper_conf_asplos_sivathanucsz19_b200/lib/libastra.so paper_conf_asplos_sivathanucsz19_b200/lib/libastra_base.so
git stash pop -q
cp /tmp/libastra_new.so paper_conf_asplos_sivathanucsz19_b200/lib/libastra.so
echo built
