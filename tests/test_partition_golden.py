"""Hand-derived pins of the sequential multi-source partition (reading R12,
Fig. 6 lines 2-8 P:156-170), for the oracle and the library."""
import pytest

import oracle
from oracle import PlanError, ERR_NO_SPACE
import paper_conf_hpca_zhouwylbyx23_b200 as mp

G = 4096
BW = [[0, 0, 1, 1], [0, 0, 1, 1], [0] * 4, [0] * 4]
SPARE = [0, 0, 10 * G, 10 * G]


def test_two_sources_one_copy_each():
    """Source 0 (6 units) plans first against 10/10 units: 3/3 (equal
    links).  Source 1 (8 units) then sees 7/7: 4/4."""
    reqs = [(1, [8 * G], 1), (0, [6 * G], 1)]          # order of the list does not matter
    part, plans = oracle.sequential_partition(4, SPARE, BW, reqs, G)
    assert part[0] == [0, 0, 3 * G, 3 * G] and part[1] == [0, 0, 4 * G, 4 * G]
    assert mp.partition_sequential(4, SPARE, BW, reqs, G) == part


def test_copies_split_the_remaining_spare():
    """Source 0 keeps 2 handles in flight: it plans against floor(10/2) = 5
    units per importer (3/3) and reserves 2 x 3 = 6 per importer; source 1
    then fits its 8 units into the 4/4 left."""
    reqs = [(0, [6 * G], 2), (1, [8 * G], 1)]
    part, _ = oracle.sequential_partition(4, SPARE, BW, reqs, G)
    assert part[0] == [0, 0, 6 * G, 6 * G] and part[1] == [0, 0, 4 * G, 4 * G]
    assert mp.partition_sequential(4, SPARE, BW, reqs, G) == part


def test_later_source_runs_out():
    """With 3 copies source 0 reserves 9/9 units; source 1's 8 units no
    longer fit in the 1/1 left: NO_SPACE (R9)."""
    reqs = [(0, [6 * G], 3), (1, [8 * G], 1)]
    with pytest.raises(PlanError) as ei:
        oracle.sequential_partition(4, SPARE, BW, reqs, G)
    assert ei.value.code == ERR_NO_SPACE
    with pytest.raises(mp.MPressError) as ei:
        mp.partition_sequential(4, SPARE, BW, reqs, G)
    assert ei.value.code == mp.ERR_NO_SPACE
