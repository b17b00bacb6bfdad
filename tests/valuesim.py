"""Definition-1 value simulator — an independent ground truth used to PIN the oracle.

Definition 1: "For a read on the host that can receive a value
from a write to the same variable on the accelerator (or vice versa), a data
mapping issue occurs if the read does not observe the write; namely, the read
fails to return the value placed by the write."

This simulator does not use the state machine at all.  Every write gets a
fresh id; OV and CV of each 8-byte word hold the id of the value they contain
(BOT = never defined, "the variable's CV has not been created and its
OV has not been explicitly initialized"); transfers copy contents (P:117,
P:121, Table I memcpy); new/delete CV make the CV content undefined.  A read
is an issue iff the side it reads does not hold the latest write; it is a use
of uninitialized memory iff the side holds no defined value at all, else a use
of stale data.

The map-clause reference counting is re-implemented here from Table I
 and OpenMP 5.1 independently of the oracle's code.
"""
from __future__ import annotations

BOT = 0  # undefined content

RH, WH, RT, WT, MAP_ENTER, MAP_EXIT, UPDATE = 0, 1, 2, 3, 8, 9, 10
BASE = 11                           # pointer tag -> base address (reading Z25)
CV_BASE = 16                        # the CV address of a mapped OV address (reading Z26)
CV_ADDR = 0x80                      # RT / WT arg bit: the address is a CV address (Z26)
TASK_BEGIN, TASK_END, SYNC = 12, 13, 14
TO, FROM, TOFROM, ALLOC, RELEASE, DELETE = 0, 1, 2, 3, 4, 5
ALWAYS = 0x10                       # map-type modifier bit (N4, reading Z21)
PRESENT = 0x20                      # map-type modifier bit: the section must already be mapped
UUM, USD, BO = 1, 2, 4


class MapError(Exception):
    pass


class ValueSim:
    """bo=True: the buffer-overflow extension: a target access to a
    word whose CV does not exist (no map entry created it, or it was deleted)
    does not reach this word's CV at all; it is reported as BO and changes
    nothing.  CV existence is tracked as a set of words here, not as a bit."""

    def __init__(self, bo: bool = False, unified: bool = False, devices: int = 1):
        """unified=True: unified memory (reading Z23): OV and CV are the same
        storage (one dict), so transfers, allocation and release change nothing."""
        self.bo = bo
        self.unified = unified
        self.alive: set[int] = set()      # words whose CV exists
        self.ov: dict[int, int] = {}
        self.cv: dict[int, int] = self.ov if unified else {}
        # several accelerators (reading Z24): one CV and one present table per
        # device; `self.cv` / `self.present` always name the current record's device
        self.devices = devices
        self.cvs = [self.cv] + [{} for _ in range(devices - 1)]
        self.presents = [[] for _ in range(devices)]
        self.latest: dict[int, int] = {}
        self.next_id = 1
        self.present: list[list[int]] = self.presents[0]  # [lo, hi, refcount, cv] byte intervals
        self.ignored = 0                  # word-ops of CV addresses no CV holds (Z26)
        self.issues: set[tuple[int, int, int]] = set()
        self.base: dict[int, int] = {}    # pointer tag -> base byte address (Z25)
        self.tag = 0                      # tag of the current target access

    # -- per-word primitive operations ---------------------------------------
    def _write(self, side, w):
        vid = self.next_id
        self.next_id += 1
        side[w] = vid
        self.latest[w] = vid

    def _read(self, side, w, idx):
        lat = self.latest.get(w)
        got = side.get(w, BOT)
        if lat is None or got != lat:
            self.issues.add((w, idx, UUM if got == BOT else USD))

    def _entry_of(self, byte):
        for ent in self.present:
            if ent[0] <= byte < ent[1]:
                return ent
        return None

    def word_op(self, name, w, idx):
        if self.bo and name in ("RT", "WT") and w not in self.alive:
            self.issues.add((w, idx, BO))
            return
        if self.bo and name in ("RT", "WT") and self.tag in self.base:
            # the access must land in the CV allocated for its pointer's
            # base; reaching another variable's CV is an overflow (the access still
            # reads / writes the CV it reached)
            if self._entry_of(self.base[self.tag]) is not self._entry_of(8 * w):
                self.issues.add((w, idx, BO))
        if name == "RH":
            self._read(self.ov, w, idx)
        elif name == "RT":
            self._read(self.cv, w, idx)
        elif name == "WH":
            self._write(self.ov, w)
        elif name == "WT":
            self._write(self.cv, w)
        elif self.unified and name in ("UPT", "UPH", "NEW", "DEL"):
            return                        # one storage: nothing moves, nothing is (de)allocated
        elif name == "UPT":   # memcpy(CV, OV)
            self.cv[w] = self.ov.get(w, BOT)
        elif name == "UPH":   # memcpy(OV, CV)
            self.ov[w] = self.cv.get(w, BOT)
        elif name in ("NEW", "DEL"):  # fresh or deleted CV holds nothing
            self.cv[w] = BOT
            if name == "NEW":
                self.alive.add(w)
            else:
                self.alive.discard(w)
        else:
            raise ValueError(name)

    @staticmethod
    def words(addr, length):
        return range(addr // 8, (addr + length - 1) // 8 + 1)

    # -- map clauses (Table I) ------------------------------------------------
    def _lookup(self, lo, hi):
        hit = None
        for ent in self.present:
            if ent[0] <= lo and hi <= ent[1]:
                hit = ent
            elif lo < ent[1] and ent[0] < hi:
                raise MapError("partial overlap")
        return hit

    def record(self, op, addr, length, arg, idx, tag=0):
        cv_addr = op in (RT, WT) and bool(arg & CV_ADDR)    # Z26: a device address
        if op in (RT, WT):
            arg &= ~CV_ADDR
        if self.devices > 1:              # Z24: the device of the record
            d = arg if op in (RT, WT) else (arg >> 6 if op in (MAP_ENTER, MAP_EXIT, UPDATE, CV_BASE) else 0)
            arg = arg & 0x3F if op in (MAP_ENTER, MAP_EXIT, UPDATE, CV_BASE) else arg
            self.cv, self.present = self.cvs[d], self.presents[d]
        always = bool(arg & ALWAYS)           # OpenMP 5.1 `always` map-type modifier (reading Z21)
        present = bool(arg & PRESENT)         # OpenMP 5.1 `present`: not mapped -> error
        arg &= ~(ALWAYS | PRESENT)
        if cv_addr:
            # the interval tree of P:269: which entry's CV holds this device address
            hit = [e for e in self.present if len(e) > 3 and e[3] is not None and e[3] <= addr < e[3] + e[1] - e[0]]
            if not hit:
                self.ignored += (addr + length - 1) // 8 - addr // 8 + 1
                return
            addr = hit[0][0] + (addr - hit[0][3])
        if op == CV_BASE:
            ent = self._entry_of(addr)
            if ent is not None:
                c = length - (addr - ent[0])            # w1 [0,48) carries the CV address
                for f in self.present:                  # one CV per device address: older
                    if f is not ent and f[3] is not None and f[3] < c + ent[1] - ent[0] and c < f[3] + f[1] - f[0]:
                        f[3] = None                     # overlapping placements are gone
                ent[3] = c
            return
        if op in (RH, WH, RT, WT):
            name = {RH: "RH", WH: "WH", RT: "RT", WT: "WT"}[op]
            self.tag = tag if op in (RT, WT) else 0
            for w in self.words(addr, length):
                self.word_op(name, w, idx)
            self.tag = 0
        elif op == BASE:
            self.base[tag] = addr
        elif op == MAP_ENTER:
            ent = self._lookup(addr, addr + length)
            if ent is None and present:
                raise MapError("present modifier on an unmapped section")
            if ent is not None:
                ent[2] += 1
                if always and arg in (TO, TOFROM):
                    for w in self.words(addr, length):
                        self.word_op("UPT", w, idx)
                return
            self.present.append([addr, addr + length, 1, None])
            for w in self.words(addr, length):
                self.word_op("NEW", w, idx)
            if arg in (TO, TOFROM):
                for w in self.words(addr, length):
                    self.word_op("UPT", w, idx)
        elif op == MAP_EXIT:
            ent = self._lookup(addr, addr + length)
            if ent is None:
                return
            ent[2] = 0 if arg == DELETE else ent[2] - 1
            if ent[2] != 0 and always and arg in (FROM, TOFROM):
                for w in self.words(addr, length):
                    self.word_op("UPH", w, idx)
            if ent[2] == 0:
                if arg in (FROM, TOFROM):
                    for w in self.words(addr, length):
                        self.word_op("UPH", w, idx)
                for w in self.words(ent[0], ent[1] - ent[0]):
                    self.word_op("DEL", w, idx)
                self.present.remove(ent)
        elif op == UPDATE:
            ent = self._lookup(addr, addr + length)
            if ent is None:
                return
            for w in self.words(addr, length):
                self.word_op("UPT" if arg == 0 else "UPH", w, idx)
        # TASK_BEGIN / TASK_END / SYNC: no data effect

    def run(self, records):
        """records: iterable of (w0, w1); returns the set of UUM/USD issues."""
        for idx, (w0, w1) in enumerate(records):
            w0 = int(w0)
            w1 = int(w1)
            self.record((w0 >> 48) & 0xFF, w0 & ((1 << 48) - 1), w1 & ((1 << 48) - 1),
                        w0 >> 56, idx, w1 >> 48)
        return self.issues

    def state_bits(self, w):
        """The 4 quantities of Table II as observed on values (for final-state pins)."""
        lat = self.latest.get(w)
        ov = self.ov.get(w, BOT)
        cv = self.cvs[0].get(w, BOT)
        ovv = lat is not None and ov == lat
        cvv = lat is not None and cv == lat
        bits = int(ovv) | (int(cvv) << 1) | (int(ov != BOT) << 2) | (int(cv != BOT) << 3)
        for d in range(1, self.devices):  # Z24: device d's CV valid / initialised at bits 2d+2, 2d+3
            c = self.cvs[d].get(w, BOT)
            bits |= (int(lat is not None and c == lat) << (2 * d + 2)) | (int(c != BOT) << (2 * d + 3))
        return bits | (int(w in self.alive) << 4 if self.bo else 0)


def schedule_issues(ops):
    """Definition-1 check of one schedule given as a list of (word_op_name, word)."""
    vs = ValueSim()
    for k, (name, w) in enumerate(ops):
        vs.word_op(name, w, k)
    return vs.issues
